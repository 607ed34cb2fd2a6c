# ncu --set full capture of one launch of kernel $K (regex on the demangled name) during a short bench
# run -> gpurun_out/$NAME.ncu-rep (SKIP = matching launches to skip first)
K=${K:?kernel regex}
NAME=${NAME:-$(echo $K | tr -c 'a-zA-Z0-9_\n' '_')}
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k "regex:$K" \
  --launch-skip ${SKIP:-0} -c ${COUNT:-1} -o gpurun_out/$NAME -f \
  python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_$NAME.log 2>&1
tail -2 gpurun_out/ncu_$NAME.log
