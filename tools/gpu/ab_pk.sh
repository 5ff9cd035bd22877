timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_fullsize.py -x -q > gpurun_out/pk_parity.log 2>&1; echo rc=$? >> gpurun_out/pk_parity.log
bash tools/gpu/ab.sh gpurun_out/ab_pk.txt 'C4 C1 C2' paper_conf_icppw_zhangczsdhay23_b200/libsssp_base3.so paper_conf_icppw_zhangczsdhay23_b200/libsssp_pk.so
