echo "--- cv none" >> gpurun_out/ab_small.txt; for c in C4 C3 C1; do timeout 600 python tools/ab.py --config $c --runs 8 --rounds 3 --param 11=1 paper_conf_icppw_zhangczsdhay23_b200/libsssp_cv.so >> gpurun_out/ab_small.txt 2>&1; done
echo "--- small none" >> gpurun_out/ab_small.txt; for c in C4 C3 C1; do timeout 600 python tools/ab.py --config $c --runs 8 --rounds 3 --param 11=1 paper_conf_icppw_zhangczsdhay23_b200/libsssp_small.so >> gpurun_out/ab_small.txt 2>&1; done
echo "--- small carveout 44" >> gpurun_out/ab_small.txt; for c in C4 C3 C1; do SSSP_CARVEOUT=44 timeout 600 python tools/ab.py --config $c --runs 8 --rounds 3 --param 11=1 paper_conf_icppw_zhangczsdhay23_b200/libsssp_small.so >> gpurun_out/ab_small.txt 2>&1; done
SSSP_CARVEOUT=44 SSSP_LIB=$PWD/paper_conf_icppw_zhangczsdhay23_b200/libsssp_small.so python -c "
import gen, paper_conf_icppw_zhangczsdhay23_b200 as s, torch
g=gen.kronecker(12,16,seed=1); G=s.Graph(g.row,g.col,g.w); G.reorder(); G.sssp(0,16); print('grid_ctas carveout44', G.stats()['grid_ctas'])" >> gpurun_out/ab_small.txt 2>&1
SSSP_LIB=$PWD/paper_conf_icppw_zhangczsdhay23_b200/libsssp_small.so python -c "
import gen, paper_conf_icppw_zhangczsdhay23_b200 as s, torch
g=gen.kronecker(12,16,seed=1); G=s.Graph(g.row,g.col,g.w); G.reorder(); G.sssp(0,16); print('grid_ctas default', G.stats()['grid_ctas'])" >> gpurun_out/ab_small.txt 2>&1
