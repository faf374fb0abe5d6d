#!/usr/bin/env bash
# Build an A/B variant of the library: bash tools/ab_build.sh NAME [nvcc flags...]
#   -> build/ab/libft_NAME.so (same flags as paper_conf_sosp_liuqc0hs0y24_b200/build.py + the extra ones)
set -e
cd "$(dirname "$0")/.."
name=$1; shift
mkdir -p build/ab/obj_$name
pids=()
for f in paper_conf_sosp_liuqc0hs0y24_b200/csrc/*.cu; do
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr \
    -Xcompiler -fPIC,-fvisibility=hidden -cudart static "$@" -Iinclude -c $f -o build/ab/obj_$name/$(basename $f).o &
  pids+=($!)
done
for p in "${pids[@]}"; do wait $p; done
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o build/ab/libft_$name.so build/ab/obj_$name/*.o
echo build/ab/libft_$name.so
