#!/bin/bash
# A/B two or more variant libraries across grid sizes, interleaved, twice:
#   GRIDS="128 256 512" bash tools/grid_ab.sh tagA tagB
for rep in 1 2; do for g in ${GRIDS:-128 256 512}; do for tag in "$@"; do
  VBENCH="--grid $g" bash tools/variants.sh run $tag | sed "s/^/$g r$rep /"
done; done; done
