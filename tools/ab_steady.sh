# A/B of prebuilt libraries on the multi-chunk steady-state leg (4 x 1 GiB of config 5): LIBS="a b"
set -e
L=paper_conf_ipps_weij11_b200/libwjindex.so
for rep in $(seq ${REPS:-1}); do
for v in $LIBS; do
  cp ablibs/lib_$v.so $L
  python bench.py --steps ${STEPS:-5} --warmup 3 --e2e-steps 0 --no-cpu-baseline > gpurun_out/abs_$v.json 2>gpurun_out/abs_$v.err
  python - $v <<'PY'
import json,sys
d=json.load(open(f"gpurun_out/abs_{sys.argv[1]}.json"))
s=d["steady_state"]
print(sys.argv[1], "config2", round(d["ms_per_step"],3), "steady ms/chunk", round(s["ms_per_chunk"],3), {k:round(v,3) for k,v in s["phases_ms_per_chunk"].items() if v})
PY
done; done
