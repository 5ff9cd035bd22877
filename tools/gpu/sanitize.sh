# usage: bash tools/gpu/sanitize.sh TOOL   (one compute-sanitizer tool per gpurun call)
T=$1
timeout 1500 compute-sanitizer --tool $T --print-limit 20 python tools/sanitize_cases.py > gpurun_out/sanitizer_$T.txt 2>&1; echo "rc=$?" >> gpurun_out/sanitizer_$T.txt
