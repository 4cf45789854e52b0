# A/B of a compile-time variant, interleaved on one box:
#   bash tools/ab_probe.sh "<DEFINE=VAL ...>" "<bench args 1>" "<bench args 2>" ...
defs=$1; shift
python tools/ab_build.py /tmp/ab_variant.so $defs > /tmp/ab_build.txt 2>&1 || { tail -20 /tmp/ab_build.txt; exit 1; }
run() { timeout 300 env $1 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --no-read-calibration $2 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('%-34s %-40s %10.2f %7.4f %8.2f us' % (sys.argv[1], sys.argv[2], d['value'], r['frac'], r['avg_launch_us']))" "$1" "$2"; }
for rep in 1 2 3; do for args in "$@"; do
  run X=default "$args"
  run HISQ_DSLASH_LIB=/tmp/ab_variant.so "$args"
done; done
