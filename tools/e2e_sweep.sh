# e2e leg sweep: host chunk count and postings format (one GPU)
for args in "--e2e-chunks 2" "--e2e-chunks 4" "--e2e-chunks 8" "--e2e-chunks 16" "--vbyte --e2e-chunks 4" "--vbyte --e2e-chunks 8"; do
  python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 3 $args > gpurun_out/sw.json 2>/dev/null
  python -c "import json,sys; d=json.load(open('gpurun_out/sw.json')); print(sys.argv[1:], round(d['ms_per_step'],2), 'e2e', round(d['e2e']['ms_per_step'],2), round(d['e2e']['value']), d['e2e']['d2h_bytes_per_step'])" $args
done
