#!/bin/bash
# variants/head: the committed (HEAD) sources built for A/B timing against the working tree
set -e
cd "$(dirname "$0")/.."
rm -rf variants/head /tmp/headsrc && mkdir -p variants/head /tmp/headsrc
git archive HEAD paper_conf_icpp_nobreiss22_b200 datagen include oracle tools tests | tar -x -C variants/head
python - <<'PY'
import sys
sys.path.insert(0, "variants/head/paper_conf_icpp_nobreiss22_b200")
import build
build.build(force=True)
PY
echo variants/head built
