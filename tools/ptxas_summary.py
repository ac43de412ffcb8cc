import re,sys
for f in sys.argv[1:]:
    s=open(f).read()
    for b in re.split(r"ptxas info\s*: Compiling entry function '",s)[1:]:
        name=b.split("'")[0]
        m=re.search(r'Used (\d+) registers',b); sp=re.search(r'(\d+) bytes stack frame, (\d+) bytes spill stores, (\d+) bytes spill loads',b)
        nm=re.sub(r'_ZN3psb\d+','',name)
        g=re.match(r'(\w+?_kernel)I((?:Li\d+E)+)',nm)
        print(g.group(1) if g else nm[:30], re.findall(r'Li(\d+)E', g.group(2)) if g else '', m.group(1), sp.groups())
