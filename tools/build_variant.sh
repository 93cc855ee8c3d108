# Build a variant of libmf_b200.so with extra nvcc defines into tools/bin/<name>.so (for A/B
# timing through MF_LIB=tools/bin/<name>.so).  Needs a normal build first (_build/*.o).
# usage: bash tools/build_variant.sh ring8_1 -DMF_RING8=1
set -e
name=$1; shift
R=$(cd "$(dirname "$0")/.." && pwd)
P=$R/paper_conf_hpdc_xietfl17_b200
mkdir -p $R/tools/bin
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC -I$R/include -I$P/csrc \
  --expt-relaxed-constexpr "$@" -c $P/csrc/mf_kernels.cu -o $R/tools/bin/$name.o
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $R/tools/bin/$name.so $R/tools/bin/$name.o \
  $P/_build/mf_api.o $P/_build/mf_comm.o -ldl
echo $R/tools/bin/$name.so
