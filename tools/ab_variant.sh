#!/bin/bash
# Build the current tree with extra nvcc flags into ab/libgriffin_<tag>.so
# usage: tools/ab_variant.sh <tag> "<nvcc flags>"
set -e
TAG=$1; FLAGS=$2
ROOT=$(cd "$(dirname "$0")/.." && pwd)
WT=/tmp/abv_$TAG
rm -rf "$WT"; mkdir -p "$WT"
cp -r "$ROOT/paper_conf_ppopp_0044ws18_b200" "$ROOT/include" "$WT/"
rm -f "$WT"/paper_conf_ppopp_0044ws18_b200/libgriffin.so "$WT"/paper_conf_ppopp_0044ws18_b200/csrc/*.o
(cd "$WT" && GRIFFIN_EXTRA_NVCC="$FLAGS" python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build(force=True)")
mkdir -p "$ROOT/ab"
cp "$WT/paper_conf_ppopp_0044ws18_b200/libgriffin.so" "$ROOT/ab/libgriffin_$TAG.so"
grep -A3 "intersect_kernelILb" "$WT/paper_conf_ppopp_0044ws18_b200/csrc/ptxas.log" | grep -E "spill" | tr '\n' ' '; echo
rm -rf "$WT"
