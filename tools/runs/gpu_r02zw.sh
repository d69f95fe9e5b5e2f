#!/bin/bash
# recon: CTA barrier right after the window copies are issued (not after row 0 lands), alone on HEAD
LIBS="tools/bin/lib_head.so tools/bin/lib_ebar.so tools/bin/lib_head.so tools/bin/lib_ebar.so tools/bin/lib_head.so tools/bin/lib_ebar.so" bash tools/ab_libs.sh
