# quick GPU check: build, gpu tests (optionally a -k filter), bench
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q ${TESTK:+-k "$TESTK"} > gpurun_out/t.log 2>&1; tail -5 gpurun_out/t.log
python bench.py --e2e-steps 0 --no-cpu-baseline --steps ${STEPS:-20} > gpurun_out/bench.json 2> gpurun_out/bench.err; python tools/bench_brief.py gpurun_out/bench.json
