# Quick health check on one B200: smoke, GPU tests, headline bench line.
set -x
F=gpurun_out/check; mkdir -p $F
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $F/smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > $F/pytest_gpu.log 2>&1
timeout 900 python bench.py > $F/bench_tdes.json 2> $F/bench_tdes.err
timeout 900 python bench.py --workload mm > $F/bench_mm.json 2> $F/bench_mm.err
tail -3 $F/pytest_gpu.log; cat $F/bench_tdes.json
