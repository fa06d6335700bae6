/* CPU study (this round): JP dependency levels of the DEGk intra graph of an R-MAT
   CSR dumped by graphgen (rp<scale>.bin = int64 row_ptr, ci<scale>.bin = int32
   col_idx).  Prints levels, per-level vertices/arcs and the greedy colour count.
   Priority = fmix32(v ^ Klo) ^ Khi with K = stream key (seed 42, tag VERTEX).
       gcc -O2 -o jp_levels jp_levels.c && ./jp_levels <scale> <k>            */
#include <stdio.h>
#include <stdlib.h>
#include <stdint.h>
#include <string.h>
static uint64_t mix64(uint64_t z){z^=z>>30;z*=0xBF58476D1CE4E5B9ULL;z^=z>>27;z*=0x94D049BB133111EBULL;z^=z>>31;return z;}
static uint32_t fmix32(uint32_t h){h^=h>>16;h*=0x85EBCA6Bu;h^=h>>13;h*=0xC2B2AE35u;h^=h>>16;return h;}
static uint32_t *pvv; 
static int cmp(const void*a,const void*b){int x=*(int*)a,y=*(int*)b; uint64_t kx=((uint64_t)pvv[x]<<32)|x, ky=((uint64_t)pvv[y]<<32)|y; return kx<ky?1:(kx>ky?-1:0);}
int main(int argc,char**argv){
  int s=atoi(argv[1]); int k=atoi(argv[2]); char f[64];
  sprintf(f,"rp%d.bin",s); FILE*F=fopen(f,"rb"); fseek(F,0,2); long nb=ftell(F); fseek(F,0,0);
  long n=nb/8-1; int64_t*rp=malloc(nb); fread(rp,1,nb,F); fclose(F);
  sprintf(f,"ci%d.bin",s); F=fopen(f,"rb"); int32_t*ci=malloc(rp[n]*4); fread(ci,4,rp[n],F); fclose(F);
  uint64_t K=mix64(mix64(42ULL^0x9E3779B97F4A7C15ULL)^((uint64_t)1<<32|0)); uint32_t lo=(uint32_t)K, hi=(uint32_t)(K>>32);
  pvv=malloc(n*4); for(long v=0;v<n;v++) pvv[v]=fmix32((uint32_t)v^lo)^hi;
  char*H=malloc(n); for(long v=0;v<n;v++) H[v]=(rp[v+1]-rp[v])>k; if(k<0) memset(H,1,n);
  int*ord=malloc(n*4); long nh=0; for(long v=0;v<n;v++) if(H[v]) ord[nh++]=v;
  qsort(ord,nh,4,cmp);
  int*lev=calloc(n,4); int*col=calloc(n,4); int maxl=0;
  char*forb=calloc(1<<20,1);
  for(long i=0;i<nh;i++){int v=ord[i]; int l=0; 
    for(long e=rp[v];e<rp[v+1];e++){int w=ci[e]; if(!H[w]) continue; uint64_t kw=((uint64_t)pvv[w]<<32)|w, kv=((uint64_t)pvv[v]<<32)|v; if(kw>kv){ if(lev[w]+1>l) l=lev[w]+1; forb[col[w]]=1;}}
    int c=1; while(forb[c]) c++; col[v]=c;
    for(long e=rp[v];e<rp[v+1];e++){int w=ci[e]; if(H[w]) forb[col[w]]=0;}
    lev[v]=l; if(l>maxl) maxl=l;}
  long*lv=calloc(maxl+1,8),*la=calloc(maxl+1,8); long*lmaxd=calloc(maxl+1,8);
  for(long v=0;v<n;v++) if(H[v]){ long d=0; for(long e=rp[v];e<rp[v+1];e++) d+=H[ci[e]]; lv[lev[v]]++; la[lev[v]]+=d; if(d>lmaxd[lev[v]]) lmaxd[lev[v]]=d;}
  int maxc=0; for(long v=0;v<n;v++) if(col[v]>maxc) maxc=col[v];
  printf("n %ld nh %ld levels %d maxcolor %d\n",n,nh,maxl+1,maxc);
  // cumulative: levels by size buckets
  long bucketsV[8]={0},bucketsL[8]={0},bucketsA[8]={0};
  for(int l=0;l<=maxl;l++){ int b=0; long x=lv[l]; while(x>=10 && b<7){x/=10;b++;} bucketsL[b]++; bucketsV[b]+=lv[l]; bucketsA[b]+=la[l]; }
  for(int b=0;b<8;b++) printf("ready 10^%d: levels %ld vertices %ld arcs %ld\n",b,bucketsL[b],bucketsV[b],bucketsA[b]);
  long ca=0,cv=0; for(int l=0;l<=maxl;l++){ca+=la[l];cv+=lv[l]; if(l<20||l%250==0) printf("L%d v %ld arcs %ld maxdeg %ld cumV %ld cumA %ld\n",l,lv[l],la[l],lmaxd[l],cv,ca);}
  // "tail": vertices at level>=L: count and induced arcs
  for(int L=50; L<=maxl; L*=2){ long tv=0,ta=0; for(long v=0;v<n;v++) if(H[v]&&lev[v]>=L){tv++; for(long e=rp[v];e<rp[v+1];e++){int w=ci[e]; if(H[w]&&lev[w]>=L) ta++;}} printf("tail L>=%d: vertices %ld induced arcs %ld\n",L,tv,ta);}
  FILE*o=fopen("lev.bin","wb"); fwrite(lev,4,n,o); fclose(o);
  return 0;}
