"""Quality report for bench.py and the tests: NMI of a result against the LFR planted partition.

Not a step of the Louvain path and not part of the product package (paper_conf_ppopp_wangllwm00z25_b200
is argument marshalling over the C ABI only); torch ops on the GPU are fine for a report.
"""


def nmi_device(labels, truth) -> float:
    """NMI of two partitions (Table 4; ref. [52] Strehl & Ghosh 2002:
    I(X;Y) / sqrt(H(X) H(Y))), computed on the device with torch ops for reporting the quality
    of a result against the LFR planted partition.  Not a step of the Louvain path; 0 clusters
    shared -> 0, both single-cluster -> 1 (same convention as the test oracle)."""
    import torch
    x = torch.as_tensor(labels).to("cuda", torch.int64).flatten()
    y = torch.as_tensor(truth).to("cuda", torch.int64).flatten()
    n = x.numel()
    if n == 0:
        return 1.0
    _, xi = torch.unique(x, return_inverse=True)
    _, yi = torch.unique(y, return_inverse=True)
    ky = int(yi.max()) + 1
    na = torch.bincount(xi).double()
    nb = torch.bincount(yi).double()
    pair, nab = torch.unique(xi * ky + yi, return_counts=True)
    a, b = pair // ky, pair % ky
    nab = nab.double()
    mi = float((nab / n * torch.log(n * nab / (na[a] * nb[b]))).sum())
    hx = float(-(na / n * torch.log(na / n)).sum())
    hy = float(-(nb / n * torch.log(nb / n)).sum())
    if hx == 0.0 or hy == 0.0:
        return 1.0 if hx == hy else 0.0
    return mi / (hx * hy) ** 0.5
