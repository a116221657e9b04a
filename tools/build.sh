#!/bin/bash
# Build libpsml.so (and the oracle) from anywhere; prints only errors/warnings and spill info.
cd "$(dirname "$0")/.." && python -m paper_conf_icpp_chenzzzz020_b200.build "$@" 2>&1 | grep -iE "error|warning|spill stores, [1-9]" | head -30
true
