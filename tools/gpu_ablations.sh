# f3 / f4 ablations: C5 RLE direct vs decompression vs plain; C4s sparse vs dense representation
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1
B="timeout 200 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu-baseline"
$B --config C5 > gpurun_out/abl_C5_plain.log 2>&1
$B --config C5 --rle on > gpurun_out/abl_C5_rle_direct.log 2>&1
$B --config C5 --rle on --rle-split decompress > gpurun_out/abl_C5_rle_decompress.log 2>&1
$B --config C5 --rle auto > gpurun_out/abl_C5_rle_auto.log 2>&1
$B --config C4s > gpurun_out/abl_C4s_sparse.log 2>&1
$B --config C4s --dense > gpurun_out/abl_C4s_dense.log 2>&1
$B --config C4b > gpurun_out/abl_C4b_sparse.log 2>&1
$B --config C4b --dense > gpurun_out/abl_C4b_dense.log 2>&1
$B --config C2 > gpurun_out/abl_C2_plain.log 2>&1
$B --config C2 --rle auto > gpurun_out/abl_C2_rle_auto.log 2>&1
