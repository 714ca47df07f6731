# A/B of library builds on C5's first windows (tools/c5_full.py, no oracle): per-kernel device ms
#   bash tools/ab_c5.sh <windows> lib1.so lib2.so ...
N=${1:?windows}; shift
for r in 1 2; do for L in "$@"; do
  RTM_LIB_PATH=$L C5_PROFILE=1 timeout 600 python tools/c5_full.py --windows $N --batch 1000 2>/dev/null | \
    python -c "import sys,json; ls=[json.loads(x) for x in sys.stdin if x.startswith('{')]; k=[x for x in ls if 'k_fold' in x]; d=[x for x in ls if 'reduce_device_s' in x]; print('$L', round(d[0]['reduce_device_s']*1e3,2), k[0] if k else '')"
done; done
