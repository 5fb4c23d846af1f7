# Round measurement on one B200 (everything lands in gpurun_out/final/; copy what is judged to profiles/).
set -x
F=gpurun_out/final; mkdir -p $F
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $F/smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $F/pytest_gpu.log 2>&1
timeout 900 python bench.py > $F/bench_tdes.json 2> $F/bench_tdes.err
for w in ${WORKLOADS:-mb mm mm_tc mix c5 mpe tdes_var nop}; do
  timeout 900 python bench.py --workload $w > $F/bench_$w.json 2> $F/bench_$w.err
done
timeout 600 python scripts/probe_life.py nop mm tdes mix mb c5 mpe > $F/life.jsonl 2> $F/life.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $F/launches_tdes.csv \
  python bench.py --prespawn --steps 3 --warmup 3 --no-naive --no-cpu --quick > $F/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master -s 3 -c 1 -o $F/tdes_full \
  python bench.py --workload tdes --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > $F/tdes_full.log 2>&1
python scripts/ncu_summary.py $F/tdes_full.ncu-rep > $F/ncu_tdes_full.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:master -s 3 -c 1 -o $F/mm_full \
  python bench.py --workload mm --prespawn --steps 1 --warmup 3 --no-naive --no-cpu --quick > $F/mm_full.log 2>&1
python scripts/ncu_summary.py $F/mm_full.ncu-rep > $F/ncu_mm_full.txt 2>&1
find gpurun_out/final -name "*.ncu-rep" -delete
timeout 600 python scripts/probe_busy.py mm tdes nop mb > $F/busy.jsonl 2>&1
timeout 300 python scripts/probe_session_overhead.py > $F/session_overhead.json 2>&1
timeout 600 python scripts/probe_runtime.py > $F/runtime.json 2>&1
ls -la $F
