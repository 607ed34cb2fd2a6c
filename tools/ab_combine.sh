python -m pytest tests -m gpu -x -q > gpurun_out/t.log 2>&1; tail -5 gpurun_out/t.log
for v in 1 0 1; do WJ_DOC_COMBINE=$v python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/b_$v.json 2>gpurun_out/b_$v.err
python - $v <<'PY'
import json,sys
d=json.load(open(f"gpurun_out/b_{sys.argv[1]}.json"))
print(sys.argv[1], round(d["ms_per_step"],3), d["config"]["stream_elems_per_gpu"], {k:round(v["ms_per_step"],3) for k,v in d["kernels"].items() if v["ms_per_step"]}, {k:round(v,3) for k,v in d["phases_ms_per_step"].items() if v})
PY
done
