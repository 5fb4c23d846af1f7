# Round-end re-measurement of the final binary (subset of gpu_final.sh): GPU suite, the headline and
# the workloads whose bodies changed last, the tdes launch list and ncu full captures.
set -x
F=gpurun_out/final2; mkdir -p $F
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $F/smoke.log 2>&1
timeout 600 python bench.py > $F/bench_tdes.json 2> $F/bench_tdes.err
timeout 1500 python -m pytest tests -m gpu -q > $F/pytest_gpu.log 2>&1
for w in ${WORKLOADS:-dct dct_noshm mix c5 mm64 mm}; do
  timeout 900 python bench.py --workload $w > $F/bench_$w.json 2> $F/bench_$w.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $F/launches_tdes.csv \
  python bench.py --prespawn --steps 3 --warmup 3 --no-naive --no-cpu --quick > $F/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master -s 3 -c 1 -o $F/tdes_full \
  python bench.py --workload tdes --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > $F/tdes_full.log 2>&1
python scripts/ncu_summary.py $F/tdes_full.ncu-rep > $F/ncu_tdes_full.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master -s 3 -c 1 -o $F/dct_full \
  python bench.py --workload dct --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > $F/dct_full.log 2>&1
python scripts/ncu_summary.py $F/dct_full.ncu-rep > $F/ncu_dct_full.txt 2>&1
find gpurun_out/final2 -name "*.ncu-rep" -delete
ls -la $F
