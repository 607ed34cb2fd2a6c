# build ablibs/lib_<name>.so with extra nvcc defines:  tools/build_variant.sh name [-DX=1 ...]
set -e
name=$1; shift
mkdir -p ablibs
NCCL_INC=$(python -c "from paper_conf_ipps_weij11_b200 import build as b; print(b.nccl_include())")
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared \
  -Xptxas -v "$@" -I "$NCCL_INC" -o ablibs/lib_$name.so paper_conf_ipps_weij11_b200/csrc/engine.cu -ldl 2> ablibs/ptxas_$name.txt
grep -A2 "k_tok_emit" ablibs/ptxas_$name.txt | grep -o "Used [0-9]* registers.*\|[0-9]* bytes spill stores" | head -2
