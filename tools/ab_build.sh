#!/bin/bash
# Build libft.so of git revision $1 into build/ab/libft_$2.so (same-box A/B timing; FT_LIB_PATH selects it).
set -e
REV=$1; NAME=$2
ROOT=$(cd "$(dirname "$0")/.." && pwd)
TMP=$(mktemp -d)
git -C "$ROOT" archive "$REV" | tar -x -C "$TMP"
(cd "$TMP" && python -m paper_conf_sosp_liuqc0hs0y24_b200.build --force > /dev/null)
mkdir -p "$ROOT/build/ab"
cp "$TMP/paper_conf_sosp_liuqc0hs0y24_b200/libft.so" "$ROOT/build/ab/libft_$NAME.so"
rm -rf "$TMP"
echo "$ROOT/build/ab/libft_$NAME.so"
