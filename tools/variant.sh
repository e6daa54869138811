#!/bin/bash
# Development A/B: build a copy of the repo under variants/<name>/ with extra nvcc flags.
#   tools/variant.sh <name> [nvcc flags...]      e.g. tools/variant.sh pf1 -DRP_PREFETCH=1
# Run a tool from the copy (its own librp.so): python variants/<name>/tools/ncu_cfg.py 5 0 8
set -e
name=$1; shift
root=$(cd "$(dirname "$0")/.." && pwd)
dst=$root/variants/$name
rm -rf "$dst"; mkdir -p "$dst"
(cd "$root" && tar cf - --exclude=./variants --exclude=./.git --exclude=./gpurun_out --exclude=./profiles \
   --exclude='*.so' --exclude=./paper_conf_icpp_arumugamrztgi17_b200/build . ) | (cd "$dst" && tar xf -)
cp "$root/oracle/liboracle.so" "$dst/oracle/" 2>/dev/null || true
cd "$dst" && RP_NVCC_EXTRA="$*" python -m paper_conf_icpp_arumugamrztgi17_b200.build --force > build.log 2>&1
echo "$dst"
