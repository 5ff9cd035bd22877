# usage: bash tools/gpu/ab.sh OUT CONFIGS LIB...   (A/B of library builds, pull phases on)
OUT=$1; CF=$2; shift 2
for c in $CF; do
  timeout 600 python tools/ab.py --config $c --runs 8 --rounds 3 --param 11=1 "$@" >> $OUT 2>&1
done
