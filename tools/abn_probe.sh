# A/B/C... of several compile-time variants, interleaved on one box:
#   bash tools/abn_probe.sh "<bench args>[|<more bench args>...]" "NAME1:DEF=V DEF2=V" "NAME2:DEF=V" ...
# ABN_TESTS (default 'multi_rhs or rhs8'): pytest -k filter run once per variant at the end
IFS='|' read -ra argsets <<< "$1"; shift
names=(default); libs=("")
for v in "$@"; do
  n=${v%%:*}; defs=${v#*:}
  python tools/ab_build.py /tmp/abn_$n.so $defs > /tmp/abn_$n.txt 2>&1 || { tail -20 /tmp/abn_$n.txt; exit 1; }
  names+=("$n"); libs+=("/tmp/abn_$n.so")
done
for rep in 1 2 3; do for args in "${argsets[@]}"; do for i in "${!names[@]}"; do
  if [ -z "${libs[$i]}" ]; then e="X=1"; else e="HISQ_DSLASH_LIB=${libs[$i]}"; fi
  timeout 300 env $e python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --no-read-calibration $args 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('%-12s %-30s %10.2f %7.4f %8.2f us' % (sys.argv[1], sys.argv[2], d['value'], r['frac'], r['avg_launch_us']))" "${names[$i]}" "$args"
done; done; done
for i in "${!names[@]}"; do
  if [ -z "${libs[$i]}" ]; then e="X=1"; else e="HISQ_DSLASH_LIB=${libs[$i]}"; fi
  echo "${names[$i]}: $(env $e timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full_size.py -q -x -k "${ABN_TESTS:-multi_rhs or rhs8}" 2>&1 | tail -1)"
done
