#!/bin/bash
# Build libdt.so in-tree (nvcc, sm_100a); prints errors only, then whether it is up to date.
cd "$(dirname "$0")/.." && python -c "from paper_conf_hpdc_wubvjd16_b200 import _build; _build.build()" 2>&1 | grep -iE "error|warning: v" | head -20
python -c "from paper_conf_hpdc_wubvjd16_b200 import _build; print('stale' if _build.needs_build() else 'built')"
