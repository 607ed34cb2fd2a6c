# A/B of prebuilt libraries (ablibs/lib_<name>.so): LIBS="a b", ENVS="VAR=val ..." applied to all
L=paper_conf_ipps_weij11_b200/libwjindex.so
cp $L /tmp/lib_orig.so
for rep in $(seq ${REPS:-1}); do
for v in $LIBS; do
  cp ablibs/lib_$v.so $L
  env $ENVS python bench.py --steps ${STEPS:-20} --warmup 3 --e2e-steps 0 --no-cpu-baseline $BENCH_ARGS > gpurun_out/ab_$v.json 2>gpurun_out/ab_$v.err
  python - $v <<'PY'
import json,sys
d=json.load(open(f"gpurun_out/ab_{sys.argv[1]}.json"))
print(sys.argv[1], round(d["ms_per_step"],3), d["config"].get("stream_elems_per_gpu"), {k:round(v["ms_per_step"],3) for k,v in d["kernels"].items() if v["ms_per_step"]}, {k:round(v,3) for k,v in d["phases_ms_per_step"].items() if v})
PY
done; done
cp /tmp/lib_orig.so $L
