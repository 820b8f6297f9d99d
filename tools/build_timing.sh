#!/bin/bash
# Debug build with in-kernel phase timers (-DFGR_TIMING) into tbuild/libfastgr.so (use FGR_LIB_PATH=...).
set -e
cd "$(dirname "$0")/.."
NI=$(python -c "import nvidia.nccl,os;print(os.path.dirname(nvidia.nccl.__path__[0]))")/nccl
mkdir -p tbuild
for f in paper_conf_date_liulzclly22_b200/csrc/*.cu; do
  b=$(basename $f .cu)
  /usr/local/cuda/bin/nvcc -DFGR_TIMING -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo \
    -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -Iinclude -I$NI/include --expt-relaxed-constexpr -c -o tbuild/$b.o $f &
done
wait
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -o tbuild/libfastgr.so tbuild/*.o \
  -L$NI/lib -l:libnccl.so.2 -Xlinker -rpath=$NI/lib
