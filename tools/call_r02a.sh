set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
python bench.py --e2e-steps 1 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err; head -c 1500 gpurun_out/bench.json
K=k_tok_emit NAME=emit bash tools/ncu_one.sh
K="k_rs_down2<unsigned int" NAME=down2 SKIP=1 bash tools/ncu_one.sh
ls -la gpurun_out/*.ncu-rep
