# A/B timing of prebuilt libraries with env settings on the GPU box.
#   SPECS="name[:VAR=val[,VAR=val]] ..." (ablibs/lib_<name>.so), REPS=2, STEPS=20
L=paper_conf_ipps_weij11_b200/libwjindex.so
cp $L /tmp/lib_orig.so
for rep in $(seq ${REPS:-2}); do
for spec in $SPECS; do
  name=${spec%%:*}; envs=""
  [ "$spec" != "$name" ] && envs=$(echo ${spec#*:} | tr ',' ' ')
  cp ablibs/lib_$name.so $L
  env $envs python bench.py --steps ${STEPS:-20} --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ab.json 2>/dev/null
  python - "$spec" <<'PY'
import json,sys
d=json.load(open("gpurun_out/ab.json"))
k=d["kernels"]; p=d["phases_ms_per_step"]
print(sys.argv[1], round(d["ms_per_step"],3), " ".join(f"{n}={k[n]['ms_per_step']:.3f}" for n in ("tokenize_count","tokenize_emit","sort_hist","sort_scatter","rle_emit")), " ".join(f"{n}={v:.3f}" for n,v in p.items() if v))
PY
done
done
cp /tmp/lib_orig.so $L
