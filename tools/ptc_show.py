import json, sys
t = open(sys.argv[1]).read()
for line in t.split('\n'):
    if '{' not in line:
        print(line); continue
    d = json.loads(line[line.index('{'):])
    for k in ('producers', 'prep', 'epilogue', 'mma'):
        print(' ', k, d[k])
    if 'trace' in d:
        print('  trace', {k: v for k, v in d['trace'].items() if k != 'first'})
        print('  first', d['trace']['first'][:16])
