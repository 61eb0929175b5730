#!/bin/bash
# Debug build with bounded spin loops recorded to host memory (-DGALLATIN_DEBUG_SPIN)
# into tools/libgallatin_dbg.so (read by tools/spin_debug.py via GALLATIN_LIB).
cd "$(dirname "$0")/.."
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC,-O2,-Wno-attributes -shared \
  -DGALLATIN_DEBUG_SPIN=20000 -Iinclude paper_conf_ppopp_mccoyp24_b200/csrc/*.cu -o tools/libgallatin_dbg.so
