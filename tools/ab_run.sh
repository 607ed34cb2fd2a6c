set -e
L=paper_conf_ipps_weij11_b200/libwjindex.so
cp ablibs/lib_${TESTLIB:-b3}.so $L
[ -n "$SKIPTEST" ] || python -m pytest tests -m gpu -x -q -k "not config2" > gpurun_out/t.log 2>&1 || true
[ -n "$SKIPTEST" ] || tail -2 gpurun_out/t.log
for v in ${VARIANTS:-old b3 b4}; do
  cp ablibs/lib_$v.so $L
  python bench.py --steps 20 --warmup 3 > gpurun_out/ab_$v.json 2>/dev/null
  python - "$v" <<'PY'
import json,sys
d=json.load(open(f"gpurun_out/ab_{sys.argv[1]}.json"))
k=d["kernels"]
print(sys.argv[1], round(d["ms_per_step"],3), "emit", round(k["tokenize_emit"]["ms_per_step"],3), "count", round(k["tokenize_count"]["ms_per_step"],3), "tok", round(d["phases_ms_per_step"]["tokenize"],3), "uniq", round(d["phases_ms_per_step"]["unique"],3))
PY
done
