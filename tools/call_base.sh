# session start: build, quick GPU tests, bench, ncu source captures of the downsweep and emit
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size" > gpurun_out/t.log 2>&1; tail -2 gpurun_out/t.log
python bench.py --e2e-steps 0 --no-cpu-baseline --steps 20 > gpurun_out/bench.json 2> gpurun_out/bench.err; python tools/bench_brief.py gpurun_out/bench.json
K='k_rs_down2<unsigned int' NAME=s3_down COUNT=1 SKIP=1 bash tools/ncu_one.sh
K='k_tok_emit' NAME=s3_emit COUNT=1 bash tools/ncu_one.sh
python tools/ncu_summary.py gpurun_out/s3_down.ncu-rep; python tools/ncu_summary.py gpurun_out/s3_emit.ncu-rep
python tools/ncu_lines.py gpurun_out/s3_down.ncu-rep 0 30 > gpurun_out/s3_down_lines.txt 2>&1
python tools/ncu_lines.py gpurun_out/s3_emit.ncu-rep 0 40 > gpurun_out/s3_emit_lines.txt 2>&1
