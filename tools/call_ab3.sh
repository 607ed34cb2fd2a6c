# A/B of library variants built here (ablibs/lib_<name>.so), GPU tests with the default build first
set -e
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -n "$TESTS" ]; then timeout 1200 python -m pytest tests -m gpu -x -q ${TESTK:+-k "$TESTK"} > gpurun_out/t_ab.log 2>&1 || true; tail -2 gpurun_out/t_ab.log; fi
LIBS="$LIBS" REPS=${REPS:-2} bash tools/ab_libs.sh
