#!/bin/bash
# Build a variant copy of the library under scratch/<name> with extra nvcc defines, e.g.
#   tools/mk_variant.sh pw2 -DEPI4_PROD_WARPS=2 -DEPI4_PF=2
set -e
cd "$(dirname "$0")/.."
name=$1; shift
rm -rf scratch/$name && mkdir -p scratch/$name
cp -r datagen include oracle paper_conf_icpp_nobreiss22_b200 tools tests scratch/$name/
rm -f scratch/$name/paper_conf_icpp_nobreiss22_b200/libepi4.so
python - "$name" "$@" <<'PY'
import sys
sys.path.insert(0, f"scratch/{sys.argv[1]}/paper_conf_icpp_nobreiss22_b200")
import build
build.build(force=True, extra=tuple(sys.argv[2:]))
PY
echo scratch/$name built
