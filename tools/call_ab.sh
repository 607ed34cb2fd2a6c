# A/B of emit variants: build libs, then bench each with hot default and off
set -e
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
bash tools/build_variant.sh base
bash tools/build_variant.sh s1 -DWJ_EMIT_SUB=1
bash tools/build_variant.sh m5 -DWJ_EMIT_MINB=5
bash tools/build_variant.sh s2 -DWJ_EMIT_SUB=2
LIBS="base s1 m5 s2" bash tools/ab_libs.sh
LIBS="base s1" BENCH_ARGS="--hot off" bash tools/ab_libs.sh
