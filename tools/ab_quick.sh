# quick A/B of env settings: SPECS="name:VAR=val,VAR=val ..." (same library), STEPS
for spec in ${SPECS:-base}; do
  name=${spec%%:*}; envs=""
  [ "$spec" != "$name" ] && envs=$(echo ${spec#*:} | tr ',' ' ')
  env $envs python bench.py --steps ${STEPS:-20} --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/q_$name.json 2>gpurun_out/q_$name.err
  python - $name <<'PY'
import json,sys
d=json.load(open(f"gpurun_out/q_{sys.argv[1]}.json"))
print(sys.argv[1], round(d["ms_per_step"],3), d["config"].get("stream_elems_per_gpu"), {k:round(v["ms_per_step"],3) for k,v in d["kernels"].items() if v["ms_per_step"]}, {k:round(v,3) for k,v in d["phases_ms_per_step"].items() if v})
PY
done
