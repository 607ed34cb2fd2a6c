set -e
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
bash tools/build_variant.sh base
bash tools/build_variant.sh noflush -DWJ_HOT_NO_FLUSH
bash tools/build_variant.sh noatom -DWJ_HOT_NO_FLUSH -DWJ_HOT_NO_ATOMIC
bash tools/build_variant.sh m5 -DWJ_EMIT_MINB=5
LIBS="base noflush noatom m5" BENCH_ARGS="--hot --steady-chunks 0" bash tools/ab_libs.sh
