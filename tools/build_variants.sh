#!/bin/bash
# Build variant libraries varlibs/lib_<name>.so that differ only in one source file's
# compile-time knobs (SRC=spectral (default) or ccsdt), for A/B measurements with
# tools/sweep_spectral.py / tools/time_ccsdt.py via BARRACUDA_LIB.
# Usage: [SRC=ccsdt] tools/build_variants.sh name1 "-DFLAG=.. -DFLAG2=.." name2 "..." ...
set -e
cd "$(dirname "$0")/.."
SRC=${SRC:-spectral}
python -c "import paper_conf_icpp_nelsonrbhhjn15_b200.build as b; b.build()" > /dev/null
mkdir -p varlibs
NV="/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr -Xcompiler -fPIC,-O2 -Iinclude -w"
OTHER=$(ls build/obj/*.o | grep -v "/$SRC.cu.o")
pids=()
while [ $# -ge 2 ]; do
  name=$1; flags=$2; shift 2
  ( mkdir -p build/var_$name && $NV $flags -c paper_conf_icpp_nelsonrbhhjn15_b200/csrc/$SRC.cu -o build/var_$name/$SRC.o \
    && $NV -gencode arch=compute_100a,code=sm_100a -shared -o varlibs/lib_$name.so build/var_$name/$SRC.o $OTHER -cudart static \
    && echo "built varlibs/lib_$name.so" ) &
  pids+=($!)
done
for p in "${pids[@]}"; do wait $p; done
