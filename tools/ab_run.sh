# A/B timing of prebuilt libraries (ablibs/lib_<name>.so) on the GPU box:
#   TESTLIB=<name> (GPU tests run with it first; SKIPTEST=1 skips), VARIANTS="a b a b"
set -e
L=paper_conf_ipps_weij11_b200/libwjindex.so
cp ablibs/lib_${TESTLIB:-new}.so $L
[ -n "$SKIPTEST" ] || python -m pytest tests -m gpu -x -q -k "not config2" > gpurun_out/t.log 2>&1 || true
[ -n "$SKIPTEST" ] || tail -2 gpurun_out/t.log
for v in ${VARIANTS:-old new}; do
  cp ablibs/lib_$v.so $L
  python bench.py --steps 20 --warmup 3 > gpurun_out/ab_$v.json 2>/dev/null
  python - "$v" <<'PY'
import json,sys
d=json.load(open(f"gpurun_out/ab_{sys.argv[1]}.json"))
k=d["kernels"]; p=d["phases_ms_per_step"]
print(sys.argv[1], round(d["ms_per_step"],3), " ".join(f"{n}={k[n]['ms_per_step']:.3f}" for n in ("tokenize_count","tokenize_emit","sort_hist","sort_scatter","rle_emit")), " ".join(f"{n}={v:.3f}" for n,v in p.items() if v))
PY
done
