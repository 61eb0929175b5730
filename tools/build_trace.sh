#!/bin/bash
# Debug build with refill-phase tracing (-DGALLATIN_TRACE) into tools/libgallatin_trace.so
# (read by tools/trace_phases.py / trace_refills.py via GALLATIN_LIB).
cd "$(dirname "$0")/.."
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo -Xcompiler -fPIC,-O2,-Wno-attributes -shared \
  -DGALLATIN_TRACE -Iinclude paper_conf_ppopp_mccoyp24_b200/csrc/*.cu -o tools/libgallatin_trace.so
