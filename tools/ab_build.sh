#!/bin/bash
# A/B the C5 bench across compile-time variants: tools/ab_build.sh "-DX=1" "-DX=2 -DY=3" ...
# rebuilds libstemroot.so with the extra nvcc defines for each variant, then runs tools/ab.sh;
# the default build is restored at the end.
for defs in "$@"; do
  SR_EXTRA_NVCC="$defs" python -c "import paper_conf_micro_chungnkk25_b200 as s; s.build(force=True)" || { echo "[$defs] BUILD FAILED"; continue; }
  echo -n "[$defs] "; bash tools/ab.sh "SR_VARIANT=1"
done
python -c "import paper_conf_micro_chungnkk25_b200 as s; s.build(force=True)"
