python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for tool in ${TOOLS:-memcheck racecheck synccheck}; do
  small=""; [ $tool = racecheck ] && small="--small"
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize.py $small > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -4 gpurun_out/sanitize_$tool.log
done
