#!/bin/bash
# Extract one kernel's SASS from libmcts.so: tools/sass_fn.sh <name-regex> > out.sass
cuobjdump -sass ${2:-paper_conf_ipps_rockis11_b200/libmcts.so} | awk -v pat="$1" '/Function : /{f = ($0 ~ pat)} f'
