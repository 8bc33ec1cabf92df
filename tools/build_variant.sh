#!/bin/bash
# Build libsweetknn.so from a git ref into variants/<name>.so (A/B timing via SKNN_LIB=...).
#   tools/build_variant.sh <ref> <name>
set -e
ref=$1; name=$2
root=$(cd "$(dirname "$0")/.." && pwd)
wt=/tmp/sknn_wt_$name
rm -rf "$wt"; git -C "$root" worktree prune
git -C "$root" worktree add -f --detach "$wt" "$ref" >/dev/null
python "$wt/paper_conf_icde_chends17_b200/buildlib.py" --force >/dev/null
mkdir -p "$root/variants"
cp "$wt/paper_conf_icde_chends17_b200/libsweetknn.so" "$root/variants/$name.so"
git -C "$root" worktree remove --force "$wt"
echo "$root/variants/$name.so"
