#!/bin/bash
# A/B with the asynchronous scatter: ring chunks per turn (CPT) and ring stages (NST)
VARIANTS=" ;-DGX_PB_CPT=2;-DGX_PB_NST=3; " bash tools/pb_variants.sh
