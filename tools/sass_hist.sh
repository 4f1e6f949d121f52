#!/bin/bash
# static SASS opcode histogram of one kernel of the built library: tools/sass_hist.sh <symbol-substring>
cuobjdump -sass "$(dirname $0)/../paper_conf_ispass_maxw23_b200/libtfhe_b200.so" 2>/dev/null | \
  awk -v k="$1" '/Function : /{f=index($0,k)>0} f' | grep -oE '^\s+/\*[0-9a-f]+\*/\s+(@!?U?P[0-9T] )?[A-Z0-9_.]+' | \
  awk '{print $NF}' | sed -E 's/^(IMAD(\.(HI|WIDE|IADD|MOV|SHL|U32))?).*/\1/; t; s/\..*//' | sort | uniq -c | sort -rn | head -${2:-25}
