set -e
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q -k "btree or multichunk or read_postings or many_new or config1 or multi or partials" > gpurun_out/t_probe.log 2>&1 || true; tail -2 gpurun_out/t_probe.log
bash tools/build_variant.sh base
bash tools/build_variant.sh smemp -DWJ_DS_SMEM_PEERS=1
bash tools/build_variant.sh ds64 -DWJ_DS_MAXREG=0
LIBS="base smemp ds64" BENCH_ARGS="--steady-chunks 0" REPS=2 bash tools/ab_libs.sh
python bench.py --e2e-steps 0 --no-cpu-baseline > gpurun_out/b_steady.json 2>/dev/null; python -c "
import json;d=json.load(open('gpurun_out/b_steady.json'));s=d['steady_state'];print('single', round(d['ms_per_step'],3), 'steady', round(s['ms_per_chunk'],3), s['kernels_ms_per_chunk'], s['phases_ms_per_chunk'])"
