# ncu --set full captures (one launch each) of the kernels in $KS (regexes), with source-line summaries
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for k in $KS; do
  n=$(echo $k | tr -c 'a-zA-Z0-9_\n' '_')
  K="$k" NAME="p_$n" SKIP=${SKIP:-0} bash tools/ncu_one.sh
  python tools/ncu_summary.py gpurun_out/p_$n.ncu-rep
  python tools/ncu_lines.py gpurun_out/p_$n.ncu-rep 0 30 > gpurun_out/p_${n}_lines.txt 2>&1
done
