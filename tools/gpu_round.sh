python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -3 gpurun_out/t.log
python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; cat gpurun_out/bench.json | head -c 3000
python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/ref.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches.csv > gpurun_out/launch_summary.txt 2>&1; head -40 gpurun_out/launch_summary.txt
K=k_tok_emit NAME=emit bash tools/ncu_one.sh
K="k_rs_down2<unsigned int" NAME=down2 SKIP=1 bash tools/ncu_one.sh
python tools/ncu_summary.py gpurun_out/emit.ncu-rep > gpurun_out/ncu_emit.txt 2>&1; python tools/ncu_summary.py gpurun_out/down2.ncu-rep > gpurun_out/ncu_down2.txt 2>&1
