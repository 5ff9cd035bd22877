for cv in none 58 100 0 30; do echo "--- carveout $cv" >> gpurun_out/ab_cv.txt; if [ $cv = none ]; then unset SSSP_CARVEOUT; else export SSSP_CARVEOUT=$cv; fi; for c in C4 C3; do timeout 600 python tools/ab.py --config $c --runs 8 --rounds 2 --param 11=1 paper_conf_icppw_zhangczsdhay23_b200/libsssp_cv.so >> gpurun_out/ab_cv.txt 2>&1; done; done
unset SSSP_CARVEOUT
