#!/bin/bash
# Instruction mix of one flux kernel instantiation's SASS (main loop = whole body).
# usage: tools/sass_stats.sh '<mangled-name-regex>'
cd "$(dirname "$0")/.."
F=$(cuobjdump -elf paper_conf_ipps_heislersdms24_b200/libbte.so 2>/dev/null | grep -o "_ZN3bte[A-Za-z0-9_]*" | sort -u | grep -E "$1" | head -1)
echo "$F" | c++filt
cuobjdump -sass -fun "$F" paper_conf_ipps_heislersdms24_b200/libbte.so 2>/dev/null | grep -E "^\s+/\*[0-9a-f]+\*/" | awk '{$NF=""; print}' > /tmp/sass_$$.txt
echo "total $(wc -l < /tmp/sass_$$.txt)  LDG $(grep -c LDG /tmp/sass_$$.txt)  STG $(grep -c STG /tmp/sass_$$.txt)  DFMA $(grep -cE 'DFMA|DMUL|DADD' /tmp/sass_$$.txt)"
awk '{print $2}' /tmp/sass_$$.txt | sed 's/\..*//;s/^@!*P[0-9T]*$//' | sort | uniq -c | sort -rn | head -14 | tr '\n' ' '; echo
rm -f /tmp/sass_$$.txt
