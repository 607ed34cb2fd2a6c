python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests -m gpu -x -q -k "hot or partials or multi" > gpurun_out/t_hot.log 2>&1; tail -2 gpurun_out/t_hot.log
for a in "" "--hot" "" "--hot"; do python bench.py --e2e-steps 0 --no-cpu-baseline $a > gpurun_out/b_hot.json 2>/dev/null; echo "args=$a"; python tools/bench_brief.py gpurun_out/b_hot.json 2>/dev/null | head -3; python -c "
import json;d=json.load(open('gpurun_out/b_hot.json'))['steady_state'];print('steady', round(d['ms_per_chunk'],3))"; done
