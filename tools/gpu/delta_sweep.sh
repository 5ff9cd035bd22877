SSSP_LIB=$PWD/paper_conf_icppw_zhangczsdhay23_b200/libsssp_cg.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "kronecker_parity or hub or pull or bf_tail or fig" > gpurun_out/cg_parity.log 2>&1; echo rc=$? >> gpurun_out/cg_parity.log
bash tools/gpu/ab.sh gpurun_out/ab_cg.txt 'C4 C3' paper_conf_icppw_zhangczsdhay23_b200/libsssp_base5.so paper_conf_icppw_zhangczsdhay23_b200/libsssp_cg.so
timeout 900 python tools/ab.py --config C4 --runs 8 --rounds 2 --param 11=1 paper_conf_icppw_zhangczsdhay23_b200/libsssp_base5.so --deltas 10 12 14 16 18 20 24 > gpurun_out/delta_sweep.txt 2>&1
timeout 900 python tools/ab.py --config C3 --runs 8 --rounds 2 --param 11=1 paper_conf_icppw_zhangczsdhay23_b200/libsssp_base5.so --deltas 0.06 0.08 0.1 0.12 0.15 >> gpurun_out/delta_sweep.txt 2>&1
timeout 900 python tools/ab.py --config C1 --runs 8 --rounds 2 --param 11=1 paper_conf_icppw_zhangczsdhay23_b200/libsssp_base5.so --deltas 32 48 64 96 128 >> gpurun_out/delta_sweep.txt 2>&1
