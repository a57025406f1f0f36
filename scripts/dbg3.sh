#!/bin/bash
P=tricore+1f,tricore+3f,tricore+6f,fig4,clique4,k4core+2f,diamondcore+2f,c4core+2f,clique5
for v in "" "FSGC_NO_VENN_TERMS=1" "FSGC_PUBLISH=0"; do env $v timeout 120 python scripts/debug_variants.py pl2k $P 2; done
for v in "" "FSGC_NO_EDGE_TERMS=1" "FSGC_PUBLISH=0"; do env $v timeout 120 python scripts/debug_variants.py rmat16x 4-tailed-triangle,3-tailed-triangle 2 2>&1 | tail -4; done
