set -x
python tools/ab_build.py /tmp/p111.so HISQ_MRHS_PIPE=1 > /tmp/b.txt 2>&1 || tail /tmp/b.txt
O=gpurun_out/r03_ncu8; mkdir -p $O
A="--steps 8 --warmup 3 --no-cpu-baseline --no-e2e --no-read-calibration --nrhs 8"
python bench.py $A > $O/plain_default.txt 2>&1 && \
  ncu --set full --clock-control none --import-source on -k regex:dslash -s 5 -c 1 -o $O/def -f python bench.py $A > $O/ncu_def.txt 2>&1
HISQ_DSLASH_LIB=/tmp/p111.so python bench.py $A > $O/plain_p111.txt 2>&1 && \
  HISQ_DSLASH_LIB=/tmp/p111.so ncu --set full --clock-control none --import-source on -k regex:dslash -s 5 -c 1 -o $O/p111 -f python bench.py $A > $O/ncu_p111.txt 2>&1
for n in def p111; do
  ncu -i $O/$n.ncu-rep --page raw --csv > $O/${n}_raw.csv 2>&1
  ncu -i $O/$n.ncu-rep --page source --csv > $O/${n}_source.csv 2>&1
  ncu -i $O/$n.ncu-rep --page details --csv > $O/${n}_details.csv 2>&1
done
ls -la $O
