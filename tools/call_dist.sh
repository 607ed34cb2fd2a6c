python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q -k "multi or stem" > gpurun_out/t_dist.log 2>&1; tail -3 gpurun_out/t_dist.log
python bench.py --e2e-steps 0 --no-cpu-baseline --steady-chunks 0 > gpurun_out/b1.json 2>/dev/null; python tools/bench_brief.py gpurun_out/b1.json | head -2
WJ_BENCH_FORCE_DIST=1 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --e2e-steps 0 --no-cpu-baseline --steady-chunks 0 > gpurun_out/bench_dist1.json 2> gpurun_out/bench_dist1.err; python tools/bench_brief.py gpurun_out/bench_dist1.json; tail -2 gpurun_out/bench_dist1.err
