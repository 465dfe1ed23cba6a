#!/bin/bash
# Build libatos.so from a git revision (default HEAD) into variants/libatos_<rev>.so for A/B timing (tools only).
set -e
REV=${1:-HEAD}
ROOT=$(cd "$(dirname "$0")/.." && pwd)
TMP=$(mktemp -d)
git -C "$ROOT" archive "$REV" paper_conf_icpp_chenbpbyo22_b200/csrc include | tar -x -C "$TMP"
mkdir -p "$ROOT/variants"
OUT="$ROOT/variants/libatos_${REV}.so"
OBJS=()
for f in "$TMP"/paper_conf_icpp_chenbpbyo22_b200/csrc/*.cu; do
  o="$TMP/$(basename "$f" .cu).o"
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC \
    -Xcompiler -fvisibility=hidden -I "$TMP/include" -I "$TMP/paper_conf_icpp_chenbpbyo22_b200/csrc" \
    --expt-relaxed-constexpr -c "$f" -o "$o" &
  OBJS+=("$o")
done
wait
/usr/local/cuda/bin/nvcc -shared -gencode arch=compute_100a,code=sm_100a -cudart static -o "$OUT" "${OBJS[@]}" -ldl -lpthread -lrt
rm -rf "$TMP"
echo "$OUT"
