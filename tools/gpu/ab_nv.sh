SSSP_LIB=$PWD/paper_conf_icppw_zhangczsdhay23_b200/libsssp_nv.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/nv_parity.log 2>&1; echo rc=$? >> gpurun_out/nv_parity.log
bash tools/gpu/ab.sh gpurun_out/ab_nv.txt 'C4 C3 C1' paper_conf_icppw_zhangczsdhay23_b200/libsssp_base4.so paper_conf_icppw_zhangczsdhay23_b200/libsssp_nv.so
