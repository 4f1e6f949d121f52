#!/bin/bash
# per-barrier-section SASS opcode histogram of one kernel: tools/sass_sections.sh <lib.so> <mangled-name-substring>
cuobjdump -sass "$1" 2>/dev/null | awk -v k="$2" '/Function : /{f=index($0,k)>0} f' | \
  awk '/BAR.SYNC|BAR.ARV|BAR.RED/{n++} {print n"\t"$0}' | grep -E '^\S+\s+/\*[0-9a-f]+\*/' | \
  awk -F'\t' '{sec=$1; split($2,a," "); op=a[2]; if(op ~ /^@/) op=a[3]; sub(/;$/,"",op); key=op; if (key !~ /^IMAD/) sub(/\..*/,"",key); c[sec" "key]++} END{for(k in c) print k, c[k]}' | \
  sort -k1,1n -k3,3nr | awk '{if($1!=p){print "--- section "$1; p=$1} if($3>=4) print "   "$2, $3}'
