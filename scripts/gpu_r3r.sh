# 2 forwarders (CE, 4 MTBs/SM): runtime tests under CE; life cycle of 3DES / MM (where the non-body time is)
F=gpurun_out/r3r; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
PAGODA_TEST_FLAGS=0x40 timeout 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_ce_ingest.py -q -k "four or ce or ring or sessions or pool or lifecycle" > $F/pytest.log 2>&1; tail -2 $F/pytest.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "mm_config3 or mm_tc or mm_noshm" > $F/pytest_mm.log 2>&1; tail -2 $F/pytest_mm.log
for i in 1 2; do timeout 200 python bench.py --workload mm --quick --no-configs 2>/dev/null | tail -1 > $F/mm_0_$i.json; done
python scripts/ab_summary.py $F > $F/ab.txt 2>&1; cat $F/ab.txt
timeout 300 python scripts/probe_life.py tdes mm > $F/life.jsonl 2> $F/life.err; cat $F/life.jsonl
