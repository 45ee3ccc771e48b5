#!/bin/bash
# A/B of compile-time variants on a few layers: bash scripts/ab_variants.sh "<flags1>" "<flags2>" ...
cd "$(dirname "$0")/.."
LAYERS=${LAYERS:-"res2a_branch2c:4 res3a_branch2c:4 res4a_branch2c:4 res2a_branch2c:8"}
for flags in "$@"; do
  python paper_conf_icpp_hanhyylhgwwlq20_b200/_build.py $flags > /dev/null 2>&1 || { echo "build failed: $flags"; continue; }
  echo "== $flags"
  python scripts/time_layer.py $LAYERS 2>&1 | grep -v Warning
done
