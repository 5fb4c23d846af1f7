# Round-end evidence pass on one B200 (run under gpurun):  OUT=final_r2b bash scripts/gpu_evidence.sh
# the GPU suite (and the runtime suites again with every context on the copy-engine ingest), smoke + its launch list,
# the default bench line (all five configs), the pool at --gpus 2, the headline's launch list, ncu --set full captures
# of the MasterKernel on four workloads (self-draining sessions).
F=gpurun_out/${OUT:-evidence}; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > $F/pytest_gpu.log 2>&1
PAGODA_TEST_FLAGS=0x40 timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_bruteforce.py tests/test_gpu_ce_ingest.py -q > $F/pytest_gpu_ce.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $F/smoke.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $F/launches_smoke.csv python -c "import __graft_entry__ as g; g.smoke()" > $F/smoke_ncu.log 2>&1
timeout 1200 python bench.py > $F/bench_default.json 2> $F/bench_default.err
timeout 600 python bench.py --gpus 2 --workload c5 --steps 5 > $F/bench_pool_c5.json 2> $F/bench_pool_c5.err
timeout 600 python bench.py --gpus 2 --steps 10 > $F/bench_pool_tdes.json 2> $F/bench_pool_tdes.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $F/launches_tdes.csv python bench.py --quick --no-configs --prespawn --steps 2 --warmup 1 > $F/launches_run.log 2>&1
# (MM on the doorbell ingest at its preset arena: a kernel profiled under ncu is serialised against the copy
#  engine's stream, so a copy-engine-ingest session cannot be captured)
for w in tdes mm mix mb; do
  X=""; [ $w = mm ] && X="--ce 0"
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:master_kernel -c 1 -o $F/ncu_$w python bench.py --workload $w --quick --no-configs --prespawn --steps 1 --warmup 0 $X > $F/ncu_${w}_run.log 2>&1
  python scripts/ncu_summary.py $F/ncu_$w.ncu-rep > $F/ncu_${w}_full.txt 2>&1
done
# (compute-sanitizer is closed on the GPU pool since round 2's first session: profiles/r2_sanitizer_*.txt are those runs)
rm -f $F/*.ncu-rep   # the summaries above are what is kept (gpurun_out merges at most 64 MiB)
tail -3 $F/pytest_gpu.log; tail -3 $F/pytest_gpu_ce.log; tail -2 $F/smoke.log; grep -c master_kernel $F/launches_smoke.csv
