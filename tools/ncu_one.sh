# ncu --set full capture of one launch of kernel $K (regex) during a short bench run -> gpurun_out/$K.ncu-rep
K=${K:?kernel regex}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -c ${COUNT:-1} -o gpurun_out/$K -f \
  python bench.py --steps 1 --warmup 1 --e2e-steps 0 --no-cpu-baseline > gpurun_out/ncu_$K.log 2>&1
tail -3 gpurun_out/ncu_$K.log
