#!/bin/bash
# usage: tools/sass_hist.sh <lib.so> <function-name-regex>  -> opcode histogram of that function
cuobjdump -sass "$1" | awk -v pat="$2" '/Function : /{p = ($0 ~ pat)} p' | grep -E "^\s+/\*[0-9a-f]{4}\*/" | sed -E 's/^\s+\/\*[0-9a-f]+\*\/\s+//; s/^@!?U?P[0-9T] //' | awk '{print $1}' | sort | uniq -c | sort -rn
