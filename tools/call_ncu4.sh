# ncu --set full captures of the postings kernels (one launch each) on config 2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for k in k_rle_write_tma k_copy_by_rank k_rle_count k_lexrank; do
  K="$k" NAME="r02_$k" bash tools/ncu_one.sh
  python tools/ncu_summary.py gpurun_out/r02_$k.ncu-rep
done
