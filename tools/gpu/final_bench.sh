# Round-end measurement set: every config's bench line, the reference (oracle) arm, the C4 launch list and
# one ncu --set full capture of the persistent kernel. Outputs under gpurun_out/final/.
mkdir -p gpurun_out/final
O=gpurun_out/final
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $O/gpu.txt
timeout 600 python bench.py > $O/bench_C4.json 2> $O/bench_C4.err; echo "C4 rc=$?" >> $O/rc.txt
for c in C1 C2 C3; do timeout 600 python bench.py --config $c > $O/bench_$c.json 2> $O/bench_$c.err; echo "$c rc=$?" >> $O/rc.txt; done
timeout 600 python bench.py --no-reorder --steps 16 > $O/bench_C4_noreorder.json 2> $O/bench_C4_noreorder.err; echo "noreorder rc=$?" >> $O/rc.txt
timeout 900 python bench.py --config C5 --multi > $O/bench_C5_multi.json 2> $O/bench_C5_multi.err; echo "C5 rc=$?" >> $O/rc.txt
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference.json 2> $O/bench_reference.err; echo "ref rc=$?" >> $O/rc.txt
timeout 300 python bench.py --profile --steps 2 --warmup 1 > $O/plain.log 2>&1 && \
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/launches_c4.csv python bench.py --profile --steps 2 --warmup 1 > $O/ncu_launch.log 2>&1 && \
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_delta_step -s 3 -c 1 -o $O/prof_c4 python bench.py --profile --steps 2 --warmup 1 > $O/ncu_full.log 2>&1
echo "ncu rc=$?" >> $O/rc.txt
