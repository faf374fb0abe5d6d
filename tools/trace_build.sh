# Build the development-only traced library libft_trace.so (role timing counters; -DFT_TRACE).
set -e
cd "$(dirname "$0")/.."
mkdir -p build/trace
for f in paper_conf_sosp_liuqc0hs0y24_b200/csrc/*.cu; do
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr \
    -Xcompiler -fPIC,-fvisibility=hidden -cudart static -DFT_TRACE $EXTRA -Iinclude -c $f -o build/trace/$(basename $f).o
done
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o build/trace/libft_trace${SUFFIX}.so build/trace/*.o
echo build/trace/libft_trace.so
