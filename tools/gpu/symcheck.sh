timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "symmetric or pull or fig" > gpurun_out/sym_parity.log 2>&1; echo rc=$? >> gpurun_out/sym_parity.log
for c in C4 C3; do timeout 300 python tools/time_symcheck.py $c; SSSP_LIB=$PWD/paper_conf_icppw_zhangczsdhay23_b200/libsssp_base5.so timeout 300 python tools/time_symcheck.py $c; done > gpurun_out/symcheck.txt 2>&1
