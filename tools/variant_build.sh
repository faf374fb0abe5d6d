#!/bin/bash
# Build the working tree's libft.so with extra nvcc flags into build/ab/libft_$1.so (same-box A/B
# timing of compile-time variants; FT_LIB_PATH selects it).  usage: tools/variant_build.sh NAME "-DFOO ..."
set -e
NAME=$1; shift
ROOT=$(cd "$(dirname "$0")/.." && pwd)
OBJ=$ROOT/build/var_$NAME; mkdir -p $OBJ $ROOT/build/ab
for f in $ROOT/paper_conf_sosp_liuqc0hs0y24_b200/csrc/*.cu; do
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr \
    -Xcompiler -fPIC,-fvisibility=hidden -cudart static $* -I$ROOT/include -c $f -o $OBJ/$(basename $f).o &
done
wait
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o $ROOT/build/ab/libft_$NAME.so $OBJ/*.o
echo $ROOT/build/ab/libft_$NAME.so
