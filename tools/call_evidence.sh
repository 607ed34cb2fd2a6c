# round evidence at HEAD on one B200 (GPU tests run separately): smoke, bench (e2e + CPU baseline), dist
# path at N=1 through torchrun, reference arm, launch list with DRAM bytes, ncu --set full of the top
# kernels, compute-sanitizer memcheck / racecheck / synccheck on a small corpus
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err; python tools/bench_brief.py gpurun_out/bench_full.json
WJ_BENCH_FORCE_DIST=1 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --e2e-steps 0 --no-cpu-baseline --steady-chunks 0 > gpurun_out/bench_dist1.json 2> gpurun_out/bench_dist1.err; python tools/bench_brief.py gpurun_out/bench_dist1.json
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/ref.json 2> gpurun_out/ref.err; head -c 300 gpurun_out/ref.json; echo
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline --steady-chunks 0 > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches.csv 1 --json gpurun_out/ncu_traffic.json --bmin 1976511937 > gpurun_out/launch_summary.txt 2>&1; head -14 gpurun_out/launch_summary.txt
for k in k_tok_emit "k_rs_down2<unsigned.long,..bool.0,..bool.0,..bool.1,..bool.0" k_rlw_write k_tok_count k_copy_by_rank; do
  n=$(echo $k | tr -c 'a-zA-Z0-9_\n' '_' | cut -c1-40)
  K="$k" NAME="e_$n" bash tools/ncu_one.sh > /dev/null 2>&1
  python tools/ncu_summary.py gpurun_out/e_$n.ncu-rep
done
python tools/trace_step.py > gpurun_out/trace_head.txt 2>/dev/null; tail -1 gpurun_out/trace_head.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/t_full.log 2>&1; tail -2 gpurun_out/t_full.log
