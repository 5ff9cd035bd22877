for c in C4 C3; do timeout 300 python tools/trace_run.py --config $c --runs 3 --param pull_symmetric=1 2>&1 | grep -v "^\s*|" | head -80; done > gpurun_out/tr_final.txt 2>&1
