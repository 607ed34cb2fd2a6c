# one gpurun call: build, GPU tests (TESTS=-k expression, or "all"), then an A/B of library variants
#   VARIANTS="name:-DX=1 name2:" (distinct names; empty defines = the default build), REPS, BENCH_ARGS (ab_libs.sh)
set -e
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -n "$TESTS" ]; then
  if [ "$TESTS" = all ]; then
    timeout 2400 python -m pytest tests -m gpu -x -q > gpurun_out/t_ab.log 2>&1 || true
  else
    timeout 2400 python -m pytest tests -m gpu -x -q -k "$TESTS" > gpurun_out/t_ab.log 2>&1 || true
  fi
  tail -3 gpurun_out/t_ab.log
fi
names=""
for v in $VARIANTS; do
  n=${v%%:*}; d=${v#*:}
  bash tools/build_variant.sh $n $(echo $d | tr ',' ' ')
  names="$names $n"
done
names="$PREBUILT $names"  # PREBUILT: ablibs/lib_<name>.so built here from another commit
[ -z "${names// }" ] || LIBS="$names" bash tools/ab_libs.sh
