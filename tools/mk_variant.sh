#!/bin/bash
# Build a variant copy of the library under variants/<name> with extra nvcc defines, e.g.
#   tools/mk_variant.sh pw2 -DEPI4_PROD_WARPS=2 -DEPI4_PF=2
set -e
cd "$(dirname "$0")/.."
name=$1; shift
rm -rf variants/$name && mkdir -p variants/$name
cp -r datagen include oracle paper_conf_icpp_nobreiss22_b200 tools tests variants/$name/
rm -f variants/$name/paper_conf_icpp_nobreiss22_b200/libepi4.so
python - "$name" "$@" <<'PY'
import sys
sys.path.insert(0, f"variants/{sys.argv[1]}/paper_conf_icpp_nobreiss22_b200")
import build
build.build(force=True, extra=tuple(sys.argv[2:]))
PY
echo variants/$name built
