python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:emit<\(bool\)1" -c 1 -o gpurun_out/emit_hot -f python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline --steady-chunks 0 --hot > gpurun_out/ncu_emit_hot.log 2>&1; tail -1 gpurun_out/ncu_emit_hot.log
bash tools/call_sanitize.sh
