#!/bin/bash
# Build libgriffin.so of another commit into ab/libgriffin_<tag>.so (for A/B probes:
# GRIFFIN_LIBRARY=ab/libgriffin_<tag>.so python tools/stage_probe.py c2).
set -e
REV=${1:?commit}
TAG=${2:-$REV}
ROOT=$(cd "$(dirname "$0")/.." && pwd)
WT=/tmp/ab_$TAG
rm -rf "$WT"
git -C "$ROOT" worktree add -f "$WT" "$REV" >/dev/null 2>&1 || { git -C "$ROOT" worktree prune; git -C "$ROOT" worktree add -f "$WT" "$REV"; }
(cd "$WT" && python -c "from paper_conf_ppopp_0044ws18_b200 import _build; _build.build()")
mkdir -p "$ROOT/ab"
cp "$WT/paper_conf_ppopp_0044ws18_b200/libgriffin.so" "$ROOT/ab/libgriffin_$TAG.so"
git -C "$ROOT" worktree remove --force "$WT"
echo "$ROOT/ab/libgriffin_$TAG.so"
