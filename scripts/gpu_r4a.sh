# the whole GPU suite with every context on the copy-engine ingest
F=gpurun_out/r4a; mkdir -p $F
python -c "import __graft_entry__ as g; g.build()" > $F/build.log 2>&1
PAGODA_TEST_FLAGS=0x40 timeout 1500 python -m pytest tests -m gpu -q > $F/pytest_all_ce.log 2>&1; tail -5 $F/pytest_all_ce.log
