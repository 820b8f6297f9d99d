#!/bin/bash
# Build build_t/libfastgr_tt.so: the library with FGR_TREE_TIMING per-phase clock64 prints in k_dp_tree
# (use with FGR_LIB_PATH=build_t/libfastgr_tt.so).  Reuses the other objects of build/.
set -e
cd "$(dirname "$0")/.."
SITE=$(python -c "import nvidia.nccl,os;print(os.path.dirname(nvidia.nccl.__path__[0]))")
mkdir -p build_t
/usr/local/cuda/bin/nvcc -DFGR_TREE_TIMING -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC \
  -Xcompiler -fvisibility=hidden -Iinclude -I$SITE/nccl/include --expt-relaxed-constexpr -c -o build_t/dp_tree.o \
  paper_conf_date_liulzclly22_b200/csrc/dp_tree.cu
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -o build_t/libfastgr_tt.so \
  $(ls build/*.o | grep -v dp_tree) build_t/dp_tree.o -L$SITE/nccl/lib -l:libnccl.so.2 -Xlinker -rpath=$SITE/nccl/lib -Xcompiler -fPIC
