set -x
SSSP_LIB=$PWD/paper_conf_icppw_zhangczsdhay23_b200/libsssp_diag.so timeout 300 python tools/trace_run.py --config C4 --runs 3 --samples > gpurun_out/trace_diag.txt 2>&1
SSSP_LIB=$PWD/paper_conf_icppw_zhangczsdhay23_b200/libsssp_lat.so timeout 300 python tools/trace_run.py --config C4 --runs 3 --samples --quiet > gpurun_out/trace_lat.txt 2>&1
timeout 300 python bench.py --profile --steps 2 --warmup 1 > gpurun_out/plain.log 2>&1 && timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_delta_step -s 3 -c 1 -o gpurun_out/prof_c4 python bench.py --profile --steps 2 --warmup 1 > gpurun_out/ncu.log 2>&1
echo done
