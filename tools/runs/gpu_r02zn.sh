#!/bin/bash
# recon period-loop unroll (on top of the per-warp tile barriers) A/B vs base
LIBS="tools/bin/lib_base.so tools/bin/lib_wbar_u2.so tools/bin/lib_base.so tools/bin/lib_wbar_u2.so tools/bin/lib_base.so tools/bin/lib_wbar_u2.so" bash tools/ab_libs.sh
