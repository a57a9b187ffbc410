# Build lib/librdm_<name>.so with extra nvcc flags for one source file (timing experiments).
#   bash tools/build_variant.sh <name> <source.cu> "<flags>"
set -e
name=$1; src=$2; flags=$3
NCCL_DIR=$(python -c "import sysconfig;print(sysconfig.get_paths()['purelib'])")/nvidia/nccl
mkdir -p build/var
base=$(basename $src .cu)
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -I$NCCL_DIR/include -Iinclude \
  --expt-relaxed-constexpr $flags -c paper_conf_ipps_kurtysps23_b200/csrc/$base.cu -o build/var/${base}_$name.o
objs=$(ls build/obj/*.o | grep -v "/$base.o")
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o paper_conf_ipps_kurtysps23_b200/lib/librdm_$name.so $objs build/var/${base}_$name.o \
  -L$NCCL_DIR/lib -l:libnccl.so.2 -Xlinker -rpath=$NCCL_DIR/lib
