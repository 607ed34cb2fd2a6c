python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
nproc; free -g | head -2
timeout 3000 python tools/fullsize_parity.py --configs 4 --out gpurun_out/fullsize_c4.json > gpurun_out/fullsize_c4.log 2>&1; tail -2 gpurun_out/fullsize_c4.log
timeout 3000 python tools/fullsize_parity.py --configs 5 --chunks 16 --no-invariants --out gpurun_out/fullsize_c5.json > gpurun_out/fullsize_c5.log 2>&1; tail -2 gpurun_out/fullsize_c5.log
