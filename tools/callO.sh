# r01j: new handle-cycle test; bin-threshold sweep (results are threshold-independent, P7)
mkdir -p gpurun_out
make -s -j8 all >/dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "handle_cycles or across_handles or graph_mode" > gpurun_out/o_pytest.txt 2>&1; echo "exit $?" >> gpurun_out/o_pytest.txt
AB='[{}, {"bin_warp":64}, {"bin_warp":96}, {"bin_warp512":256}, {"bin_warp512":384}, {"bin_sub32":24}, {"bin_sub16":12}, {"block_split":512}, {"block_split":2048}]'
for C in lfr1m orkut rmat_lj; do echo "== $C" >> gpurun_out/o_ab_bins.txt; timeout 600 python tools/ab.py $C "$AB" >> gpurun_out/o_ab_bins.txt 2>&1; done
