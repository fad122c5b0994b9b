"""Top source lines of one kernel in an ncu report by warp-stall samples
(ncu -i REP --page source --print-source=cuda,sass), with the dominant stall reasons."""
import collections
import csv
import io
import subprocess
import sys


def main(rep, kernel_regex=None, top=25, fn_sub=None):
    args = ['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source=cuda,sass']
    if kernel_regex:
        args += ['-k', 'regex:' + kernel_regex]
    out = subprocess.check_output(args, text=True, stderr=subprocess.DEVNULL)
    per = collections.defaultdict(lambda: [0, collections.Counter(), '', 0])
    fname = ''
    hdr = None
    total = 0
    itotal = [0]
    keep = True
    for row in csv.reader(io.StringIO(out)):
        if not row:
            continue
        if row[0] == 'Function Name':
            keep = fn_sub is None or fn_sub in row[1]
            continue
        if not keep:
            continue
        if row[0] == 'File Path':
            fname = row[1].split('/')[-1]
            continue
        if row[0] == 'Line No':
            hdr = row
            continue
        if hdr is None or len(row) < len(hdr) or not row[0].isdigit():
            continue
        try:
            s = int(row[hdr.index('Warp Stall Sampling (All Samples)')] or 0)
        except ValueError:
            continue
        try:
            ins = int(row[hdr.index('Instructions Executed')] or 0)
        except ValueError:
            ins = 0
        if s == 0 and ins == 0:
            continue
        key = (fname, int(row[0]))
        per[key][3] += ins
        itotal[0] += ins
        per[key][0] += s
        per[key][2] = row[1][:70]
        total += s
        for i, h in enumerate(hdr):
            if h.startswith('stall_') and row[i] not in ('', '0'):
                try:
                    per[key][1][h[6:]] += int(float(row[i]))
                except ValueError:
                    pass
    print(f'total samples {total}, warp instructions {itotal[0]}')
    for (f, ln), (s, st, src, ins) in sorted(per.items(), key=lambda x: -x[1][0])[:top]:
        reasons = ' '.join(f'{k}:{v}' for k, v in st.most_common(2))
        print(f'{100 * s / max(total, 1):5.1f}% inst {100 * ins / max(itotal[0], 1):5.1f}% {f}:{ln:<5d} {src:60s} {reasons}')


if __name__ == '__main__':
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None, int(sys.argv[3]) if len(sys.argv) > 3 else 25,
         sys.argv[4] if len(sys.argv) > 4 else None)
