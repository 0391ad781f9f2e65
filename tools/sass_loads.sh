#!/bin/bash
# usage: tools/sass_loads.sh <object> <regex-of-mangled-name>  -> compressed LDG/FFMA/LDS sequence
obj=$1; pat=$2
for f in $(cuobjdump -sass $obj | grep Function | awk '{print $3}' | grep -E "$pat"); do
  echo "== $f"
  cuobjdump -sass -fun "$f" $obj 2>/dev/null | grep -E "^\s+/\*[0-9a-f]+\*/" | awk '{print $2}' | grep -E "^(LDG|FFMA|LDS|IMAD|STG|SHFL|BAR|@)" | sed -E 's/\..*//' | uniq -c | tr -s ' ' | tr '\n' ' ' | head -c 700; echo
done
