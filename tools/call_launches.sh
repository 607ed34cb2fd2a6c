# launch list with DRAM bytes of one config-2 index pass (ncu, serialised cold-cache) + its summary
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
[ -z "$TESTK" ] || { timeout 1200 python -m pytest tests -m gpu -x -q -k "$TESTK" > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log; }
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline --steady-chunks 0 > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches.csv 1 --json gpurun_out/ncu_traffic.json --bmin 1976511937 > gpurun_out/launch_summary.txt 2>&1; head -40 gpurun_out/launch_summary.txt
