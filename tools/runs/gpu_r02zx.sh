#!/bin/bash
# fused res-block strip height: 240 (HEAD: 3 strips per 720p frame, 288 CTAs per 16-job launch) vs 180 (384) vs 144 (480)
LIBS="tools/bin/lib_head.so tools/bin/lib_rb180.so tools/bin/lib_rb144.so tools/bin/lib_head.so tools/bin/lib_rb180.so tools/bin/lib_rb144.so" bash tools/ab_libs.sh
